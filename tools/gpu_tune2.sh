python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 900 python tools/tune.py C2 reps=2 "" "server_combine=6" "server_workers=5" "publish=0" "ro_streak=4" "ro_streak=16" "client_warps=368" "ro_adaptive=0" 2>&1 | cut -c1-200
timeout 600 python bench.py --no-cpu-baseline | tail -1 | cut -c1-300
