set -x
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "fused_step or c4_full_size_step or c2_full_size_100 or invalid or c1_all or edge_cases" 2>&1 | tail -4 > gpurun_out/s13_pytest_quick.txt
for r in 1 2 3; do
  for v in prev new; do
    case $v in prev) L=$PWD/build/libigk_prev.so;; new) L=;; esac
    IGK_LIB=$L timeout 300 python bench.py --steps 100 --no-cpu-baseline --no-repartition > gpurun_out/s13_c2_${v}_$r.json 2>/dev/null
  done
done
for v in prev new; do
  case $v in prev) L=$PWD/build/libigk_prev.so;; new) L=;; esac
  IGK_LIB=$L timeout 300 python bench.py --config C4 --steps 15 --no-cpu-baseline --no-repartition > gpurun_out/s13_c4_${v}.json 2>/dev/null
done
IGK_DEBUG_PHASES=1 timeout 300 python tools/phase_profile.py 30 C2 > gpurun_out/s13_phase_c2.txt 2>&1
cat gpurun_out/s13_pytest_quick.txt
