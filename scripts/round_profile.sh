#!/bin/bash
# One GPU session: bench (default workload), ncu launch list, per-launch DRAM
# traffic, and a full ncu capture of the contraction kernel.  Outputs in gpurun_out/.
set -x
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:pask_ -c 400 --csv \
    --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
for m in resnet50 mobilenet_v2 bert_base_fa; do
  n=$(python -c "from workloads import build_model; print(len(build_model('$m')[0]['layers']))")
  ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum -k regex:pask_ \
      -s $n -c $n --csv --log-file gpurun_out/dram_$m.csv python bench.py --model $m --steps 2 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
  python scripts/dram_traffic.py gpurun_out/dram_$m.csv $m
done
cp profiles/dram_traffic.json gpurun_out/dram_traffic.json
PASK_LINEINFO=1 python -c "from paper_conf_dac_huangdxz25_b200 import build; build.build(force=True)" > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:pask_conv_igemm -s 80 -c 3 \
    -o gpurun_out/igemm_full -f python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:pask_attention -s 14 -c 1 \
    -o gpurun_out/attention_full -f python bench.py --model bert_base_fa --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_full_attn.log 2>&1
