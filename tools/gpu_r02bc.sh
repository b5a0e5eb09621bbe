# round-2 call bc: G32 predict tree-block size sweep around 48 MB
D=gpurun_out/r02bc; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
for b in 41943040 50331648 58720256 44040192 50331648 41943040; do
  PEXP_CASES=env BF_PREDICT_BLOCK_BYTES=$b timeout 600 python tools/predict_exp.py 200 10000000 2>&1 | grep -v "^trees" | sed "s/^/blk=$b /" | head -2
done
