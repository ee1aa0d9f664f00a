python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "gsrb or fused or chunk or decomposition or c3 or vcycle or fcycle or solve" 2>&1 | grep -E "^E|passed|failed" | head -8
for n in 128 256 512; do python scripts/prof_gsrb.py $n 4 fused; done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for n in 256 512; do
  timeout 300 ncu --metrics $M --clock-control none -k regex:gsrb_pair -s 2 -c 1 --csv python scripts/prof_gsrb.py $n 3 fused 2>/dev/null | grep -E '"(dram__|gpu__)' | awk -F'","' -v c="n=$n" '{print c, $(NF-2), $(NF-1), $NF}'
done
