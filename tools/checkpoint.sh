#!/bin/bash
# Full measurement pass on the GPU box (run under gpurun): GPU tests, bench (both arms), launch lists
# (cfg 2 bench step, cfg 4 step), one ncu --set full capture of the dominant kernels.
# usage: tools/checkpoint.sh TAG
tag=$1
o=gpurun_out/ck_$tag
mkdir -p $o
timeout 900 python -m pytest tests -m gpu -q > $o/pytest_gpu.log 2>&1; tail -2 $o/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $o/smoke.log 2>&1; tail -1 $o/smoke.log
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 1 --steps 5 --warmup 3 --no-compare --no-cpu-baseline > $o/bench_torchrun1.json 2> $o/bench_torchrun1.err; tail -c 300 $o/bench_torchrun1.json
timeout 900 python bench.py > $o/bench.json 2> $o/bench.err; tail -c 600 $o/bench.json
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $o/bench_ref.json 2> $o/bench_ref.err; tail -c 300 $o/bench_ref.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file $o/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-compare --no-cpu-baseline --t-sweep "" --workloads "" --t-sweep-vgg11 "" > /dev/null 2>&1
python tools/launches.py $o/launches.csv > $o/launches.txt 2>&1; head -30 $o/launches.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file $o/launches_cfg4.csv \
    python tools/prof_step.py --workload cfg4_resnet_dvs --steps 1 > /dev/null 2>&1
python tools/launches.py $o/launches_cfg4.csv > $o/launches_cfg4.txt 2>&1; head -20 $o/launches_cfg4.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file $o/launches_cfg3.csv \
    python tools/prof_step.py --workload cfg3_vgg11 --steps 1 > /dev/null 2>&1
python tools/launches.py $o/launches_cfg3.csv > $o/launches_cfg3.txt 2>&1; head -20 $o/launches_cfg3.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"conv_lif_kernel|gemm_tc_kernel|layer0_fwd|lif_bwd_kernel" -s 30 -c 8 \
    -o $o/full python tools/prof_step.py --steps 2 > $o/ncu_full.log 2>&1; tail -2 $o/ncu_full.log
