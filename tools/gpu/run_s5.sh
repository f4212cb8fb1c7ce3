set -x
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -5 > gpurun_out/s5_pytest.txt
timeout 400 python bench.py --config C4 --steps 15 --cpu-iters 2 --no-repartition > gpurun_out/s5_bench_c4.json 2> gpurun_out/s5_bench_c4.err
timeout 300 python tools/phase_profile.py 8 C4 > gpurun_out/s5_phase_c4.txt 2>&1
for k in 2 8 32 64; do for f in 0.001 0.003 0.01 0.03 0.1; do
  timeout 200 python bench.py --config C3 --k $k --frac $f --steps 20 --no-cpu-baseline --no-repartition > gpurun_out/s5_c3_k${k}_f${f}.json 2>/dev/null
done; done
cat gpurun_out/s5_pytest.txt
