P=paper_conf_ipps_maggionibl13_b200
for rep in 1 2; do
for lib in libcme.so libcme_nobackoff.so libcme_backoff256.so; do
CME_LIBRARY=$PWD/$P/$lib timeout 600 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 CME_VI=1 2>&1 | grep "^\[" | sed "s/^/$lib /"
done; done
