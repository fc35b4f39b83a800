for cfg in "block_threads=256" "block_threads=128 max_threads=75776" "block_threads=128 max_threads=85248" "block_threads=128 max_threads=94720" "block_threads=128 max_threads=104192" "block_threads=64 max_threads=85248"; do
  python tools/one_launch.py --config bank --mode hv --launches 4 --set $cfg | tail -1 | cut -c1-60 | sed "s/^/[$cfg] /"; done
