#!/bin/bash
# quick bench on the GPU box: value, ms/step and per-class kernel times (no cpu baseline / sweeps)
# usage: tools/qb.sh TAG [extra bench.py args]
tag=$1; shift
python bench.py --steps 20 --warmup 5 --no-compare --no-cpu-baseline --t-sweep "" --workloads "" --t-sweep-vgg11 "" "$@" > gpurun_out/qb_$tag.json 2> gpurun_out/qb_$tag.err
python -c "
import json,sys
d=json.loads(open('gpurun_out/qb_$tag.json').read().strip().splitlines()[-1])
print('$tag', round(d['value'],1), round(d['ms_per_step'],3), d.get('kernels'), d['roofline']['frac'])
"
