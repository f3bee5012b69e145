#!/bin/bash
# One GPU session: bench (default workload) + reference arm, ncu launch list,
# per-launch DRAM traffic per model, and full ncu captures of the contraction
# and attention kernels.  Outputs in gpurun_out/ prefixed with $R (default r02).
set -x
R=${R:-r03}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${R}_build.log 2>&1
python bench.py > gpurun_out/${R}_bench.json 2> gpurun_out/${R}_bench.err
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${R}_bench_reference.json 2> gpurun_out/${R}_bench_reference.err
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:pask_ -c 400 --csv \
    --log-file gpurun_out/${R}_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --cold-samples 0 > /dev/null 2>&1
for m in resnet50 mobilenet_v2 bert_base_fa; do
  n=$(python -c "from workloads import build_model; print(len(build_model('$m')[0]['layers']))")
  ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum -k regex:pask_ \
      -s $n -c $n --csv --log-file gpurun_out/${R}_dram_$m.csv python bench.py --model $m --steps 2 --warmup 1 \
      --no-cpu-baseline --cold-samples 0 > /dev/null 2>&1
  python scripts/dram_traffic.py gpurun_out/${R}_dram_$m.csv $m
done
cp profiles/dram_traffic.json gpurun_out/${R}_dram_traffic.json
PASK_LINEINFO=1 python -c "from paper_conf_dac_huangdxz25_b200 import build; build.build(force=True)" > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:pask_conv_igemm -s 80 -c 3 \
    -o gpurun_out/${R}_igemm_full -f python bench.py --steps 2 --warmup 1 --no-cpu-baseline --cold-samples 0 \
    > gpurun_out/${R}_ncu_full.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:pask_attention -s 14 -c 1 \
    -o gpurun_out/${R}_attention_full -f python bench.py --model bert_base_fa --steps 2 --warmup 1 --no-cpu-baseline \
    --cold-samples 0 > gpurun_out/${R}_ncu_full_attn.log 2>&1
python -c "from paper_conf_dac_huangdxz25_b200 import build; build.build(force=True)" > /dev/null 2>&1
python scripts/trace_inference.py resnet50 > gpurun_out/${R}_trace_resnet50.log 2>&1
python scripts/trace_inference.py resnet50 --clock > gpurun_out/${R}_trace_clock_resnet50.log 2>&1
