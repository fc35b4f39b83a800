#!/usr/bin/env bash
# Refresh the round's sweep profiles (run under gpurun; outputs in gpurun_out/).
#   bash tools/refresh_profiles.sh r02 [bench] [fig5] [eb] [scaling]
tag=${1:-r02}; shift
what=${*:-"bench fig5 eb scaling"}
mkdir -p gpurun_out
for w in $what; do
  case $w in
    bench) timeout 900 python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err; echo "bench rc=$?";;
    fig5) timeout 900 python tools/fig5.py --out gpurun_out/${tag}_fig5.jsonl > gpurun_out/${tag}_fig5.log 2>&1; echo "fig5 rc=$?";;
    eb) timeout 1500 python tools/eb_sweep.py --out gpurun_out/${tag}_eb_sweep.jsonl > /dev/null 2> gpurun_out/${tag}_eb_sweep.err; echo "eb rc=$?";;
    scaling) timeout 2400 python tools/scaling_sweep.py --out gpurun_out/${tag}_scaling.jsonl > /dev/null 2> gpurun_out/${tag}_scaling.err; echo "scaling rc=$?";;
  esac
done
