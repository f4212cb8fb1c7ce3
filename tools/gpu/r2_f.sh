set -x
timeout 400 python bench.py --steps 30 --no-cpu-baseline --no-repartition > gpurun_out/f_bench_c2.json 2> gpurun_out/f_bench_c2.err
timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/f_bench_c4.json 2> gpurun_out/f_bench_c4.err
timeout 1700 python -m pytest tests -m gpu -q -x -p no:cacheprovider --durations=15 > gpurun_out/f_pytest.txt 2>&1
tail -22 gpurun_out/f_pytest.txt
