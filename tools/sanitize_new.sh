#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over the round-2 opt-in paths: the fused dgrad + reverse
# scan (conv_lif BWD, forced on at a small size) and the cross-segment weight gradients; and the default
# VGG-5 path (layer 0's suspend-wait producers).  logs under gpurun_out/san2/.  usage: tools/sanitize_new.sh
mkdir -p gpurun_out/san2
run() {  # tag env... -- cfg
  local tag=$1; shift
  for tool in memcheck racecheck synccheck; do
    log=gpurun_out/san2/${tool}_${tag}.log
    env "$@" timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/san_step.py $CFG > $log 2>&1
    echo "$tool $tag ($CFG) rc=$? : $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' $log | tr '\n' ' ') $(grep -E 'loss' $log | tail -1)"
  done
}
CFG="vgg5 14 3 2 skip" run bwd_fusion_pair SKIPPER_BWD_FUSION=1 SKIPPER_CL_MIN_UNITS=0
CFG="vgg5 14 3 2 skip" run bwd_fusion_single SKIPPER_BWD_FUSION=1 SKIPPER_CL_MIN_UNITS=0 SKIPPER_CL_PAIR=0
CFG="tiny_conv 24 3 4 skip" run wgrad_overlap SKIPPER_WGRAD_OVERLAP=1
CFG="vgg5 14 2 2 skip" run vgg5_default SKIPPER_NONE=0
