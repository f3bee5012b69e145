#!/bin/bash
# Round-2 evidence session (one GPU): ncu launch list, per-launch DRAM traffic,
# full ncu captures of the contraction kernel (L2 flushed by ncu and L2 warm),
# the persistent-tile kernel at batch 128 (tensor pipe), the scheme comparison
# (Baseline / PaSK / PaSK-I / PaSK-R / Ideal, n = 20 fresh processes per
# config) and the Table II batch sweep.  Outputs gpurun_out/${R}_*.
R=${R:-r2p}
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${R}_build.log 2>&1
B="--no-cpu-baseline --cold-samples 0 --no-configs --py-cold-samples 0"
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:pask_ -c 400 --csv \
    --log-file gpurun_out/${R}_launches.csv python bench.py --steps 2 --warmup 1 $B > /dev/null 2>&1
for m in resnet50 mobilenet_v2 bert_base_fa; do
  n=$(python -c "from workloads import build_model; print(len(build_model('$m')[0]['layers']))")
  ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum -k regex:pask_ \
      -s $n -c $n --csv --log-file gpurun_out/${R}_dram_$m.csv python bench.py --model $m --steps 2 --warmup 1 \
      $B > /dev/null 2>&1
  python scripts/dram_traffic.py gpurun_out/${R}_dram_$m.csv $m
done
cp profiles/dram_traffic.json gpurun_out/${R}_dram_traffic.json
PASK_LINEINFO=1 python -c "from paper_conf_dac_huangdxz25_b200 import build; build.build(force=True)" > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:pask_conv_igemm -s 80 -c 3 \
    -o gpurun_out/${R}_igemm_full -f python bench.py --steps 2 --warmup 1 $B > gpurun_out/${R}_ncu_full.log 2>&1
ncu --set full --clock-control none --cache-control none --import-source on -k regex:pask_conv_igemm -s 80 -c 3 \
    -o gpurun_out/${R}_igemm_full_l2warm -f python bench.py --steps 2 --warmup 1 $B > gpurun_out/${R}_ncu_full_warm.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:pask_conv_igemm_pt -s 8 -c 4 \
    -o gpurun_out/${R}_igemm_pt_b128_full -f python bench.py --batch 128 --steps 2 --warmup 1 $B \
    > gpurun_out/${R}_ncu_pt.log 2>&1
python -c "from paper_conf_dac_huangdxz25_b200 import build; build.build(force=True)" > /dev/null 2>&1
for m in resnet50 mobilenet_v2 tiny_cnn bert_base; do
  timeout 1500 python scripts/cold_samples.py --model $m --n 20 > gpurun_out/${R}_schemes_$m.log 2>&1
done
for b in 1 4 16 64 128; do
  timeout 900 python bench.py --batch $b --steps 30 --warmup 5 --no-configs --py-cold-samples 0 --cold-samples 10 \
      --timeline-samples 3 > gpurun_out/${R}_bench_batch$b.json 2> gpurun_out/${R}_bench_batch$b.err
done
