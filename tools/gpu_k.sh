# filter hash count A/B on the locked single-CTA bank worker (16-bit slots)
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
for k in 3 2 4; do
CSMV_NVCC_EXTRA="-DCSMV_BANK_FILT_K=$k" python paper_conf_ipps_nunesc022_b200/build.py --force > /dev/null
timeout 300 python tools/tune.py C2 reps=2 "server_workers=6" 2>&1 | sed "s/^/k=$k /" | cut -c1-230
done
