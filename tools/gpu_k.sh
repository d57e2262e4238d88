# filter hash count A/B on the locked single-CTA bank worker
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
P="timeout 120 python tools/probe.py"
B="C2 n_tx=16777216 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=8 ro_adaptive=1"
show() { python -c "import json,sys
for l in sys.stdin:
  d=json.loads(l); print('$1', round(d['tx_per_s']/1e6,1), 'M', round(d['abort_rate'],4), {k:v['update'] for k,v in d['aborts'].items()}, round(d['server_lock_cycles']/d['batches']))"; }
$P $B reps=2 | show k3
CSMV_NVCC_EXTRA="-DCSMV_BANK_FILT_K=2" python paper_conf_ipps_nunesc022_b200/build.py --force > /dev/null
$P $B reps=2 | show k2
$P $B server_workers=5 reps=1 | show k2w5
CSMV_NVCC_EXTRA="-DCSMV_BANK_FILT_K=1" python paper_conf_ipps_nunesc022_b200/build.py --force > /dev/null
$P $B reps=2 | show k1
