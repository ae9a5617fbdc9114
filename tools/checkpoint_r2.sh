#!/bin/bash
# Round-2 measurement pass on the GPU box (run under gpurun): GPU tests + smoke, the default bench line (both
# arms, torchrun N=1), launch lists of cfg 2/3/4 SKIP steps, per-class ncu evidence of cfg 2 and cfg 4 steps,
# one ncu --set full capture of the dominant kernel's launches.  usage: tools/checkpoint_r2.sh TAG
tag=$1
o=gpurun_out/ck_$tag
mkdir -p $o
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $o/pytest_gpu.log 2>&1; tail -2 $o/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $o/smoke.log 2>&1; tail -1 $o/smoke.log
timeout 1200 python bench.py --steps 20 --warmup 5 > $o/bench.json 2> $o/bench.err; tail -c 400 $o/bench.json
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 1 --steps 20 --warmup 5 --no-compare --no-cpu-baseline > $o/bench_torchrun1.json 2> $o/bench_torchrun1.err; tail -c 200 $o/bench_torchrun1.json
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $o/bench_ref.json 2> $o/bench_ref.err; tail -c 300 $o/bench_ref.json
for w in cfg2_vgg5 cfg3_vgg11 cfg4_resnet_dvs; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off -c 4000 --csv --log-file $o/launches_$w.csv \
      python tools/ncu_classes.py run --workload $w --out $o/launchrec_$w > /dev/null 2>&1
  python tools/launches.py $o/launches_$w.csv > $o/launches_$w.txt 2>&1; head -12 $o/launches_$w.txt
done
bash tools/ncu_classes.sh cfg2_vgg5 cfg2_$tag
bash tools/ncu_classes.sh cfg4_resnet_dvs cfg4_$tag
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"conv_lif_kernel" -s 40 -c 6 \
    -o $o/full_conv_lif python tools/prof_step.py --steps 2 > $o/ncu_full.log 2>&1; tail -1 $o/ncu_full.log
