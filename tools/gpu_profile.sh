#!/bin/bash
# One documented GPU-box runner (run through gpurun from the repo root):
#   gpurun --timeout 3000 -- 'bash tools/gpu_profile.sh TAG [STEP...]'
# Steps (default: all):
#   roofs   tools/ubench/roofs.cu + filt16_ubench.cu    -> gpurun_out/TAG/roofs.json, filt16.txt
#   tests   pytest -m gpu                               -> gpurun_out/TAG/pytest_gpu.log
#   bench   bench.py C2/C3/C4 lines (cpu_baseline on)   -> gpurun_out/TAG/bench_{c2,c3,c4}.json
#   launch  ncu launch list of the C2 bench command     -> gpurun_out/TAG/launches_c2.csv
#   ncu     ncu --set full of one timed step per config -> gpurun_out/TAG/ncu_{c2,c3,c4}.{ncu-rep,raw.csv}
#   san     compute-sanitizer memcheck/synccheck, C1    -> gpurun_out/TAG/sanitizer_*.log
# Everything is bounded by its own timeout (no step may hang the box).
set -u
TAG=${1:?tag}
shift
STEPS=${*:-roofs tests bench launch ncu san}
OUT=gpurun_out/$TAG
mkdir -p "$OUT"
NVCC="nvcc -gencode arch=compute_100a,code=sm_100a -O3"
python -c "from paper_conf_ipps_nunesc022_b200 import build; build.build()" || exit 1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv > "$OUT/nvidia_smi.txt"
NCU_M="dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum,sm__sass_inst_executed_op_shared_atom.sum"
for s in $STEPS; do
  case $s in
  roofs)
    (cd tools/ubench && $NVCC -o roofs roofs.cu && $NVCC -o filt16_ubench filt16_ubench.cu) &&
      timeout 120 tools/ubench/roofs > "$OUT/roofs.json" &&
      timeout 120 tools/ubench/filt16_ubench > "$OUT/filt16.txt"
    ;;
  tests)
    timeout 1500 python -m pytest tests -m gpu -q > "$OUT/pytest_gpu.log" 2>&1
    tail -3 "$OUT/pytest_gpu.log"
    ;;
  bench)
    for c in C2 C3 C4; do
      timeout 600 python bench.py --config $c --steps 5 --warmup 3 > "$OUT/bench_${c,,}.json" 2> "$OUT/bench_${c,,}.err"
      head -c 300 "$OUT/bench_${c,,}.json"; echo
    done
    ;;
  launch)
    timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
      --log-file "$OUT/launches_c2.csv" python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
    ;;
  ncu)
    for c in C2 C3 C4; do
      # the 4th csmv_fused launch = the first timed step (3 warm-ups), L2 flushed before it
      timeout 1200 ncu --set full --metrics "$NCU_M" --import-source on --clock-control none \
        -k regex:csmv_fused -s 3 -c 1 -f -o "$OUT/ncu_${c,,}" \
        python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline > "$OUT/ncu_${c,,}.log" 2>&1
      ncu -i "$OUT/ncu_${c,,}.ncu-rep" --page raw --csv > "$OUT/ncu_${c,,}.raw.csv" 2>/dev/null
      ncu -i "$OUT/ncu_${c,,}.ncu-rep" --page details > "$OUT/ncu_${c,,}.details.txt" 2>/dev/null
    done
    ;;
  san)
    for tool in memcheck synccheck racecheck; do
      timeout 900 compute-sanitizer --tool $tool --print-limit 20 python -c "
import sys; sys.path.insert(0, '.')
from paper_conf_ipps_nunesc022_b200 import csmv, workloads
cfg = workloads.c1(n_tx=2222, log_mode=0, watchdog_ms=600000)
with csmv.Store(cfg.n_items, cfg.n_versions) as st:
    st.load(cfg.init_values()); s = st.run(cfg.workload, cfg.n_tx, cfg.seed)
    print('committed', s['committed'], 'aborts', s['total_aborts'])
" > "$OUT/sanitizer_$tool.log" 2>&1
      tail -2 "$OUT/sanitizer_$tool.log"
    done
    ;;
  esac
done
ls "$OUT"
