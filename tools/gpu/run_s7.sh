set -x
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -5 > gpurun_out/s7_pytest.txt
for r in 1 2 3; do
  IGK_LIB=$PWD/build/libigk_head.so timeout 300 python bench.py --steps 100 --no-cpu-baseline --no-repartition > gpurun_out/s7_c2_head_$r.json 2>/dev/null
  timeout 300 python bench.py --steps 100 --no-cpu-baseline --no-repartition > gpurun_out/s7_c2_new_$r.json 2>/dev/null
done
timeout 400 python bench.py --config C4 --steps 15 --no-cpu-baseline --no-repartition > gpurun_out/s7_bench_c4.json 2>/dev/null
IGK_LIB=$PWD/build/libigk_head.so timeout 400 python bench.py --config C4 --steps 15 --no-cpu-baseline --no-repartition > gpurun_out/s7_bench_c4_head.json 2>/dev/null
timeout 300 python tools/phase_profile.py 8 C4 > gpurun_out/s7_phase_c4.txt 2>&1
timeout 200 python bench.py --config C3 --k 64 --frac 0.1 --steps 20 --no-cpu-baseline --no-repartition > gpurun_out/s7_c3_k64_f0.1.json 2>/dev/null
timeout 200 python bench.py --config C5 --steps 15 --no-cpu-baseline --no-repartition > gpurun_out/s7_bench_c5.json 2>/dev/null
cat gpurun_out/s7_pytest.txt
