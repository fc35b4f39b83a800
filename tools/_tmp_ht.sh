for i in 1 2; do for d in 0 1; do for m in hv tbv; do python tools/one_launch.py --config ht_c2 --mode $m --launches 3 --set lock_log_at_commit=$d | tail -1 | cut -c1-60 | sed "s/^/[defer=$d] /"; done; done; done
python tools/one_launch.py --config bank --mode hv --launches 3 | tail -1 | cut -c1-60
timeout 600 python -m pytest tests -m gpu -q -x -k "pipelined_at_most or lock_log_at_commit or livelock" 2>&1 | tail -1
