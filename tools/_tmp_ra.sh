for m in hv tbv fgl; do python tools/one_launch.py --config ra_paper --mode $m --launches 2 | tail -1 | cut -c1-70 | sed "s/^/[local] /"; done
GSTM_DEFINES="-DGSTM_SMEM_LOGS=1" python -m paper_conf_cgo_xuwglgq14_b200.build --force > /dev/null 2>&1
for m in hv tbv; do python tools/one_launch.py --config ra_paper --mode $m --launches 2 | tail -1 | cut -c1-70 | sed "s/^/[smem] /"; done
for m in hv; do python tools/one_launch.py --config bank --mode $m --launches 3 | tail -1 | cut -c1-70 | sed "s/^/[smem] /"; done
