# per-launch host times of the cold inference (PASK_DEBUG_COLD), ResNet-50, bench config (packaging 3, branches)
P=${P:-d}
python -c "import __graft_entry__ as g; g.build()" || exit 1
python -c "
import sys; sys.path.insert(0,'scripts'); sys.path.insert(0,'.')
import cold_samples as cs
print(cs.write_image('resnet50', '/tmp/r50.pmodel'))
print(cs.cfg_arg(dict(packaging=3, branches=1)))
" > gpurun_out/${P}_img.txt
CFG=$(tail -1 gpurun_out/${P}_img.txt)
for i in 1 2 3 4 5 6; do
  PASK_DEBUG_COLD=1 ./paper_conf_dac_huangdxz25_b200/pask_cold /tmp/r50.pmodel --cfg "$CFG" --device 0 >> gpurun_out/${P}_debugcold.log 2>&1
  echo --- >> gpurun_out/${P}_debugcold.log
done
tail -5 gpurun_out/${P}_debugcold.log
