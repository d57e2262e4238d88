# A/B of the spin-wait back-offs (build-time knobs in kernel.cuh)
for V in "" "-DCSMV_SLEEP_RESP=16 -DCSMV_SLEEP_PUB=8 -DCSMV_SLEEP_QUEUE=16" "-DCSMV_SLEEP_RESP=0 -DCSMV_SLEEP_PUB=0 -DCSMV_SLEEP_QUEUE=0" "-DCSMV_SLEEP_RESP=128 -DCSMV_SLEEP_QUEUE=128"; do
  echo "== variant: [$V]"
  CSMV_NVCC_EXTRA="$V" python paper_conf_ipps_nunesc022_b200/build.py --force > /dev/null || exit 1
  timeout 300 python tools/tune.py C2 reps=2 "" 2>&1 | cut -c1-90
  timeout 300 python tools/tune.py C3 reps=2 "server_recv=1,server_workers=7,server_combine=2,publish=0" 2>&1 | cut -c1-110
  timeout 300 python tools/tune.py C4 reps=2 "ro_streak=32" 2>&1 | cut -c1-90
done
