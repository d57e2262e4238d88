python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 900 python tools/tune.py C4 reps=1 "ro_streak=32" "ro_streak=32,client_warps=588" "ro_streak=32,client_warps=882" "ro_streak=32,client_warps=1176" "ro_streak=64,client_warps=1176" 2>&1 | cut -c1-160
timeout 900 python tools/tune.py C3 reps=1 "server_workers=7,server_recv=1,n_tx=4194304,client_warps=147" "server_workers=7,server_recv=1,n_tx=4194304,client_warps=588" "server_workers=7,server_recv=1,n_tx=4194304,ro_streak=32" 2>&1 | cut -c1-160
