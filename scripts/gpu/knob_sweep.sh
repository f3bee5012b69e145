# hot-path knob sweep (tuning.h experiment switches), 2 rounds, one box
P=${P:-k}
python -c "import __graft_entry__ as g; g.build()" || exit 1
for r in 1 2; do
  for sw in "" "PASK_FINE_CTAS=48" "PASK_FINE_CTAS=74" "PASK_FINE_CTAS=100" "PASK_FINE_MAXK=4096" \
            "PASK_FINE_MAXK=4096 PASK_FINE_CTAS=74" "PASK_SPLIT_FILL=1" "PASK_SPLIT_MINKB=4" \
            "PASK_FINE_CTAS=74 PASK_SPLIT_FILL=1"; do
    for m in ${MODELS:-bert_base}; do
      env $sw timeout 300 python scripts/hot_probe.py $m --steps 300 >> gpurun_out/${P}_sweep.log 2>&1
    done
  done
done
grep hot gpurun_out/${P}_sweep.log
