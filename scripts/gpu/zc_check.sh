P=${P:-z}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_modes.py -q -x > gpurun_out/${P}_pytest_modes.log 2>&1; tail -3 gpurun_out/${P}_pytest_modes.log
timeout 900 python bench.py --no-configs --cold-samples 10 --timeline-samples 5 --ablation-samples 3 --py-cold-samples 2 > gpurun_out/${P}_bench.json 2> gpurun_out/${P}_bench.err; python -c "
import json; d=json.loads([l for l in open('gpurun_out/${P}_bench.json') if l.startswith('{')][-1]); print(d['value'], d['ms_per_step'], d['e2e'], d['hot_direct_ms'])"
