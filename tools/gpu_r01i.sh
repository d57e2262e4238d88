# device KV preload: parity, full GPU suite, bench lines
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 600 python -m pytest tests/test_gpu_kv.py -q -k preload > gpurun_out/pytest_preload.log 2>&1; tail -3 gpurun_out/pytest_preload.log
timeout 300 python bench.py --config C4 --no-cpu-baseline > gpurun_out/bench_C4_r01i.json 2> gpurun_out/bench_C4_r01i.err; tail -1 gpurun_out/bench_C4_r01i.json | cut -c1-600
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_C2_r01i.json 2> gpurun_out/bench_C2_r01i.err; tail -1 gpurun_out/bench_C2_r01i.json | cut -c1-400
