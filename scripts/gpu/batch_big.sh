P=${P:-bb}
python -c "import __graft_entry__ as g; g.build()" || exit 1
for b in 64 128; do
  timeout 600 python bench.py --batch $b --steps 30 --warmup 5 --no-configs --py-cold-samples 0 --cold-samples 5 \
      --timeline-samples 2 --ablation-samples 0 --no-cpu-baseline > gpurun_out/${P}_bench_batch$b.json 2> gpurun_out/${P}_bench_batch$b.err
  tail -c 300 gpurun_out/${P}_bench_batch$b.err
done
