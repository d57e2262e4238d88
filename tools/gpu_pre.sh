python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
python tools/preload_time.py
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_preload.csv python tools/preload_time.py > /dev/null 2>&1
python - <<'P'
import csv
rows=[r for r in csv.reader(open('gpurun_out/launches_preload.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); vi=h.index('Metric Value')
for r in rows[1:30]: print(r[ki][:60], r[vi])
P
