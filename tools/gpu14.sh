python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --section WarpStateStats --section SourceCounters --import-source on --clock-control none --warp-sampling-interval 0 --warp-sampling-buffer-size 536870912 -k regex:csmv_fused -c 1 -o gpurun_out/prof_srv python tools/probe.py C2 n_tx=1048576 client_warps=294 publish=1 server_workers=8 ro_streak=8 server_combine=4 2>&1 | tail -3
