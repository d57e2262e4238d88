python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 900 ncu --section WarpStateStats --section SourceCounters --import-source on --clock-control none -k regex:csmv_fused -c 1 -o gpurun_out/prof_src python tools/probe.py C2 n_tx=4194304 client_warps=294 publish=1 server_workers=6 server_combine=8 ro_streak=8 ro_adaptive=1 log_mode=0 > gpurun_out/prof_src.log 2>&1
tail -2 gpurun_out/prof_src.log | cut -c1-200
