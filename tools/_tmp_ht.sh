for i in 1; do for m in hv tbv; do python tools/one_launch.py --config ht_c2 --mode $m --launches 3 | tail -1 | cut -c1-60 | sed "s/^/[inline] /"; done; done
GSTM_DEFINES="-DGSTM_PV_ATTR=__noinline__" python -m paper_conf_cgo_xuwglgq14_b200.build --force > /dev/null 2>&1
for i in 1; do for m in hv tbv; do python tools/one_launch.py --config ht_c2 --mode $m --launches 3 | tail -1 | cut -c1-60 | sed "s/^/[noinline] /"; done; done
python tools/one_launch.py --config eb_c3_h26_a16 --mode hv --launches 2 | tail -1 | cut -c1-60 | sed "s/^/[noinline] /"
python tools/one_launch.py --config bank --mode hv --launches 3 | tail -1 | cut -c1-60 | sed "s/^/[noinline] /"
