python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
B="C2 n_tx=16777216 publish=1 server_workers=6 ro_streak=8 ro_adaptive=1 log_mode=0"
for a in "client_warps=294 server_combine=4" "client_warps=294 server_combine=8" "client_warps=441 server_combine=8" "client_warps=588 server_combine=8" ; do timeout 120 python tools/phases.py $B $a | cut -c 150-720; done
