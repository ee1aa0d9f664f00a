# NEXT-1 DRAM evidence: ncu DRAM bytes of one 512^3 smooth (2 RB pairs) as one
# two-pair pass vs two colour-fused pairs (scripts/next1_once.py)
mkdir -p gpurun_out/next1
for k in 4 2; do
  timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sector_hit_rate.pct \
     --clock-control none --csv --log-file gpurun_out/next1/smooth_kind$k.csv python scripts/next1_once.py 512 $k > /dev/null 2>&1
  python scripts/launch_summary.py gpurun_out/next1/smooth_kind$k.csv
done
