python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
(cd alt_old && python -c "from paper_conf_ipps_nunesc022_b200 import build; build.build(force=True)") || exit 1
for i in 1 2; do
timeout 300 python tools/tune.py C2 reps=2 "server_workers=6,n_tx=16777216" 2>&1 | cut -c1-120
(cd alt_old && timeout 300 python tools/tune.py C2 reps=2 "server_workers=6,server_combine=8,ro_adaptive=1,log_mode=0,n_tx=16777216" 2>&1 | cut -c1-120)
done
