# round 2, session AJ: k_recount3 with L2 prefetch of the next tile (pairs of adjacent tiles) vs main
set -x
mkdir -p gpurun_out
AB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab
for rep in 1 2; do
for v in main l2pf; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  for c in C4 C5 C2; do env $L timeout 300 python tools/recount_ab.py $c 9 v3 >> gpurun_out/aj_rc_$v.txt 2>&1; done
done
done
IGK_LIB=$AB/libigk_l2pf.so timeout 900 python -m pytest tests/test_gpu_store.py tests/test_gpu_paths.py -q -x -p no:cacheprovider > gpurun_out/aj_pytest_l2pf.txt 2>&1
tail -2 gpurun_out/aj_pytest_l2pf.txt
for v in main l2pf; do echo "== $v"; grep -h '"ms"' gpurun_out/aj_rc_$v.txt | cut -c1-60; done
