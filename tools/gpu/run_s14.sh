set -x
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "fused_step or c4_full_size_step or c2_full_size_100 or invalid or c1_all or edge_cases or hub" 2>&1 | tail -4 > gpurun_out/s14_pytest_quick.txt
for r in 1 2 3; do
  for v in prev mid new; do
    case $v in prev) L=$PWD/build/libigk_prev.so;; mid) L=$PWD/build/libigk_mid.so;; new) L=;; esac
    IGK_LIB=$L timeout 300 python bench.py --steps 100 --no-cpu-baseline --no-repartition > gpurun_out/s14_c2_${v}_$r.json 2>/dev/null
  done
done
for v in prev mid new; do
  case $v in prev) L=$PWD/build/libigk_prev.so;; mid) L=$PWD/build/libigk_mid.so;; new) L=;; esac
  IGK_LIB=$L timeout 300 python bench.py --config C4 --steps 15 --no-cpu-baseline --no-repartition > gpurun_out/s14_c4_${v}.json 2>/dev/null
  IGK_LIB=$L timeout 300 python bench.py --config C5 --steps 15 --no-cpu-baseline --no-repartition > gpurun_out/s14_c5_${v}.json 2>/dev/null
done
cat gpurun_out/s14_pytest_quick.txt
