set -x
timeout 600 python -m pytest tests/test_shard.py -q -x -p no:cacheprovider -k "p2p" > gpurun_out/k_pytest_p2p.txt 2>&1
tail -n 30 gpurun_out/k_pytest_p2p.txt
