set -x
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -4 > gpurun_out/s8_pytest.txt
for r in 1 2 3; do
  for v in head new v_noeager v_novdch; do
    case $v in head) L=$PWD/build/libigk_head.so;; new) L=;; *) L=$PWD/build/$v/libigk.so;; esac
    IGK_LIB=$L timeout 300 python bench.py --steps 100 --no-cpu-baseline --no-repartition > gpurun_out/s8_c2_${v}_$r.json 2>/dev/null
  done
done
for v in head new v_noeager v_novdch; do
  case $v in head) L=$PWD/build/libigk_head.so;; new) L=;; *) L=$PWD/build/$v/libigk.so;; esac
  IGK_LIB=$L timeout 300 python bench.py --config C4 --steps 15 --no-cpu-baseline --no-repartition > gpurun_out/s8_c4_${v}.json 2>/dev/null
done
cat gpurun_out/s8_pytest.txt
