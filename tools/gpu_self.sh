python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 900 python tools/tune.py C2 reps=2 "server_workers=7" "server_workers=6,debug_flags=64" 2>&1 | cut -c1-150
timeout 300 python tools/tune.py C3 reps=1 "server_workers=7,n_tx=4194304" "server_workers=6,debug_flags=64,n_tx=4194304" 2>&1 | cut -c1-150
timeout 300 python tools/phases.py C2 n_tx=16777216 publish=1 server_workers=6 server_combine=8 ro_streak=8 ro_adaptive=1 log_mode=0 debug_flags=64 client_warps=294 | cut -c150-800
