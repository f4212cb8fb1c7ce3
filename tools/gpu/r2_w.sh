# round 2, session W: recount3 residual peel vs not, 256-vertex tiles (2 CTAs/SM); C2 refine arrivals with sub-phase stamps (flushed L2)
set -x
mkdir -p gpurun_out
AB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab
for rep in 1 2; do
for v in main nopeel v8m2; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  for c in C4 C5 C2; do env $L timeout 300 python tools/recount_ab.py $c 9 v3 >> gpurun_out/w_rc_$v.txt 2>&1; done
done
done
IGK_FLUSH=1 IGK_DEBUG_ARRIVALS=1 timeout 300 python tools/phase_profile.py 12 C2 > gpurun_out/w_phase_c2.txt 2>&1
for v in main nopeel v8m2; do echo "== $v"; grep -h '"ms"' gpurun_out/w_rc_$v.txt | cut -c1-60; done
