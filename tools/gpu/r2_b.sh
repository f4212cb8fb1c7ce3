# round 2, session B: per-phase roofline legs on C2-C5 + ncu of the C4 refine
set -x
timeout 400 python bench.py --steps 20 --no-cpu-baseline --no-repartition > gpurun_out/b_bench_c2.json 2> gpurun_out/b_bench_c2.err
timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/b_bench_c4.json 2> gpurun_out/b_bench_c4.err
timeout 400 python bench.py --config C5 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/b_bench_c5.json 2> gpurun_out/b_bench_c5.err
timeout 300 python bench.py --config C3 --k 64 --frac 0.1 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/b_bench_c3.json 2> gpurun_out/b_bench_c3.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_refine" -s 5 -c 1 -o gpurun_out/b_refine_c4 python tools/profile_step.py C4 5 > gpurun_out/b_ncu.log 2>&1
ls -la gpurun_out/
