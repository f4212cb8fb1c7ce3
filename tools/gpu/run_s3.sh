set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
nproc; lscpu | grep "Model name"
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/s3_pytest.txt
timeout 400 python bench.py > gpurun_out/s3_bench_c2.json 2> gpurun_out/s3_bench_c2.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s3_launches_c2.csv python bench.py --steps 3 --warmup 3 --profile > gpurun_out/s3_ncu_bench.log 2>&1
timeout 400 python bench.py --config C4 --steps 15 --cpu-iters 4 > gpurun_out/s3_bench_c4.json 2> gpurun_out/s3_bench_c4.err
cat gpurun_out/s3_pytest.txt; tail -c 800 gpurun_out/s3_bench_c2.json
