set -x
for L in build_ab/libcme_prev.so paper_conf_ipps_maggionibl13_b200/libcme.so build_ab/libcme_inline.so build_ab/libcme_prev.so paper_conf_ipps_maggionibl13_b200/libcme.so build_ab/libcme_inline.so; do
  CME_LIBRARY=$PWD/$L timeout 600 python tools/kbench.py --config cfg3a_schnakenberg_2m --blocks 10 CME_TMA=1 2>&1 | tail -1
done
for L in build_ab/libcme_prev.so paper_conf_ipps_maggionibl13_b200/libcme.so build_ab/libcme_inline.so; do
  CME_LIBRARY=$PWD/$L timeout 600 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 CME_TMA=1 2>&1 | tail -1
done
