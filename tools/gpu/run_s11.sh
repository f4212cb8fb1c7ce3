set -x
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/s11_pytest.txt
for r in 1 2 3; do
  for v in prev new; do
    case $v in prev) L=$PWD/build/libigk_prev.so;; new) L=;; esac
    IGK_LIB=$L timeout 300 python bench.py --steps 100 --no-cpu-baseline --no-repartition > gpurun_out/s11_c2_${v}_$r.json 2>/dev/null
  done
done
for v in prev new; do
  case $v in prev) L=$PWD/build/libigk_prev.so;; new) L=;; esac
  IGK_LIB=$L timeout 300 python bench.py --config C4 --steps 15 --no-cpu-baseline --no-repartition > gpurun_out/s11_c4_${v}.json 2>/dev/null
  IGK_LIB=$L timeout 300 python bench.py --config C5 --steps 15 --no-cpu-baseline --no-repartition > gpurun_out/s11_c5_${v}.json 2>/dev/null
done
cat gpurun_out/s11_pytest.txt
