set -x
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -5 > gpurun_out/s6_pytest.txt
timeout 400 python bench.py --config C4 --steps 15 --cpu-iters 2 --no-repartition > gpurun_out/s6_bench_c4.json 2> gpurun_out/s6_bench_c4.err
IGK_SPLIT_B=100000000 timeout 400 python bench.py --config C4 --steps 15 --no-cpu-baseline --no-repartition > gpurun_out/s6_bench_c4_fused.json 2> /dev/null
timeout 300 python bench.py --steps 50 --cpu-iters 20 --no-repartition > gpurun_out/s6_bench_c2.json 2> gpurun_out/s6_bench_c2.err
timeout 300 python tools/phase_profile.py 8 C4 > gpurun_out/s6_phase_c4.txt 2>&1
timeout 300 python bench.py --config C5 --steps 15 --no-cpu-baseline --no-repartition > gpurun_out/s6_bench_c5.json 2>/dev/null
for k in 2 64; do for f in 0.03 0.1; do
  timeout 200 python bench.py --config C3 --k $k --frac $f --steps 20 --no-cpu-baseline --no-repartition > gpurun_out/s6_c3_k${k}_f${f}.json 2>/dev/null
  IGK_SPLIT_B=100000000 timeout 200 python bench.py --config C3 --k $k --frac $f --steps 20 --no-cpu-baseline --no-repartition > gpurun_out/s6_c3_k${k}_f${f}_fused.json 2>/dev/null
done; done
cat gpurun_out/s6_pytest.txt
