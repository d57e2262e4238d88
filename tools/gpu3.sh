set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:csmv_fused -c 1 -o gpurun_out/prof_c2_64w python tools/probe.py C2 n_tx=262144 client_warps=64 publish=1 2>&1 | tail -5
