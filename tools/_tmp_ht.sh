python tools/one_launch.py --config ht_c2 --mode hv --launches 3 --paired 2>&1 | tail -3 | cut -c1-150
for i in 1 2; do for m in hv tbv; do python tools/one_launch.py --config ht_c2 --mode $m --launches 3 | tail -1 | cut -c1-70 | sed "s/^/[split] /"; done; done
python tools/one_launch.py --config bank --mode hv --launches 3 | tail -1 | cut -c1-70
