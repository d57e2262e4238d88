python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:csmv_fused -c 1 -o gpurun_out/prof_c2_16w python tools/probe.py C2 n_tx=131072 client_warps=16 publish=1 server_workers=4 2>&1 | tail -3
