#!/usr/bin/env bash
# One GPU pass (run under gpurun): the bench line, the roof probe, the GPU
# test suite.  Outputs land in gpurun_out/ with the given tag.
#   bash tools/gpu_check.sh r02x [bench|probe|tests ...]
tag=${1:-run}; shift
what=${*:-"bench probe tests"}
mkdir -p gpurun_out
for w in $what; do
  case $w in
    bench) timeout 900 python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err; echo "bench rc=$?";;
    probe) python tools/roof_probe.py --out gpurun_out/${tag}_roof_probe.jsonl > /dev/null 2>&1; echo "probe rc=$?";;
    tests) timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -3;;
    smoke) python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2;;
  esac
done
