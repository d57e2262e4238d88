python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
B="C2 n_tx=16777216 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=8 ro_adaptive=1"
timeout 120 python tools/phases.py $B
timeout 120 python tools/phases.py $B ro_adaptive=0
timeout 120 python tools/phases.py $B p_update_ppm=100000
timeout 120 python tools/phases.py $B p_update_ppm=0
timeout 120 python tools/phases.py $B client_warps=147
