#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over small training steps of every layer kind
# (VERDICT r1 item 10); logs under gpurun_out/san/, summary on stdout.  usage: tools/sanitize.sh
mkdir -p gpurun_out/san
for cfg in "fc784 20 4 2 skip" "tiny_fc 12 3 2 full" "tiny_conv 12 3 2 skip" "tiny_conv 12 3 2 full" "tiny_resnet 16 3 2 skip" "vgg5 14 2 2 skip"; do
  set -- $cfg
  for tool in memcheck racecheck synccheck; do
    log=gpurun_out/san/${tool}_$1_$5.log
    timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/san_step.py $cfg > $log 2>&1
    echo "$tool $cfg rc=$? : $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|LEAK SUMMARY' $log | tr '\n' ' ') $(grep -E 'loss' $log | tail -1)"
  done
done
