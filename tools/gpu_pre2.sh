python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
python tools/preload_time.py
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python bench.py --config C4 --no-cpu-baseline > gpurun_out/bench_C4_r01i.json 2> gpurun_out/bench_C4_r01i.err; tail -1 gpurun_out/bench_C4_r01i.json | cut -c1-300
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_preload.csv python tools/preload_time.py > /dev/null 2>&1
python - <<'P'
import csv
rows=[r for r in csv.reader(open('gpurun_out/launches_preload.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); vi=h.index('Metric Value')
for r in rows[1:8]: print(r[ki][:60], r[vi])
P
