set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 300 compute-sanitizer --tool memcheck --show-backtrace device python tools/probe.py C2 n_tx=65536 n_items=65536 server=1 cluster_size=2 client_warps=64 publish=1 server_workers=5 server_combine=4 ro_streak=8 2>&1 | head -40
timeout 600 ncu --set full --import-source on --clock-control none -k regex:csmv_fused -c 1 -o gpurun_out/prof_ring python tools/probe.py C2 n_tx=4194304 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=8 ro_adaptive=1 > gpurun_out/prof_ring.log 2>&1
tail -3 gpurun_out/prof_ring.log
