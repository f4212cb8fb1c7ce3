set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/g_pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g_smoke.txt 2>&1
timeout 400 python bench.py > gpurun_out/g_bench_c2.json 2> gpurun_out/g_bench_c2.err
timeout 500 python bench.py --config C4 --steps 15 --cpu-iters 3 > gpurun_out/g_bench_c4.json 2> gpurun_out/g_bench_c4.err
timeout 400 python bench.py --config C5 --steps 15 --cpu-iters 3 --no-repartition > gpurun_out/g_bench_c5.json 2> /dev/null
timeout 300 python bench.py --config C3 --k 64 --frac 0.1 --steps 20 --cpu-iters 10 --no-repartition > gpurun_out/g_bench_c3.json 2> /dev/null
timeout 300 python bench.py --config C1 --steps 15 --warmup 3 --no-repartition > gpurun_out/g_bench_c1.json 2> /dev/null
timeout 300 python tools/recount_ab.py C4 > gpurun_out/g_recount_c4.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_recount -c 1 -o gpurun_out/g_recount_c4 -f python tools/profile_run.py C4 3 --recount > /dev/null 2>&1
timeout 120 ncu -i gpurun_out/g_recount_c4.ncu-rep --page raw --csv > gpurun_out/g_recount_raw.csv 2>&1
cat gpurun_out/g_pytest.txt gpurun_out/g_smoke.txt
