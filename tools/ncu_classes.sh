#!/bin/bash
# per-class ncu evidence of one training step (tools/ncu_classes.py); usage: tools/ncu_classes.sh WORKLOAD TAG
w=$1; tag=$2; o=gpurun_out/ncu_${tag}
mkdir -p gpurun_out
timeout 1500 ncu --metrics $(python tools/ncu_classes.py metrics) --clock-control none --profile-from-start off \
    -o $o python tools/ncu_classes.py run --workload $w --out $o > $o.log 2>&1; tail -2 $o.log
python tools/ncu_classes.py summarise $o.ncu-rep ${o}_records.json > gpurun_out/ncu_${tag}.md 2>&1; head -30 gpurun_out/ncu_${tag}.md
