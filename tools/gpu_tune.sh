# build, GPU tests, then a tuning sweep (args: tune.py sets)
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 900 python tools/tune.py "$@" 2>&1
