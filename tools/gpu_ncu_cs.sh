# ncu source-level capture of the fused kernel on a reduced C2 run (server CS hotspots)
set -x
python -c "import __graft_entry__ as g; g.build()" || exit 1
TAG=${TAG:-cs}
timeout 900 ncu --set full --import-source on --clock-control none -k regex:csmv_fused -c 1 \
  -o gpurun_out/prof_$TAG python tools/probe.py C2 n_tx=4194304 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=8 ro_adaptive=1 > gpurun_out/prof_$TAG.log 2>&1
tail -3 gpurun_out/prof_$TAG.log
