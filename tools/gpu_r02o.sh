# round-2 call o: predict slots x tree-block size sweep (200-tree C4 forest, 10M query rows)
D=gpurun_out/r02o; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
for V in "BF_PREDICT_SLOTS=8" "BF_PREDICT_SLOTS=6" "BF_PREDICT_SLOTS=6 BF_PREDICT_BLOCK_BYTES=25165824" "BF_PREDICT_SLOTS=12 BF_PREDICT_BLOCK_BYTES=67108864" "BF_PREDICT_SLOTS=8 BF_PREDICT_BLOCK_BYTES=50331648" "BF_PREDICT_SLOTS=12"; do
  env $V timeout 900 python bench.py --ntree 200 --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-profile > $D/b.log 2>&1
  echo "== $V"; grep "^{" $D/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['phases_ms']['predict'],1), d['predictions_per_s'])"
done
