#!/bin/bash
# A/B of the split row layout on the products-shaped batch gather (ncu, one batch, cold L2)
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum
for S in 1 0; do
  WG_FEAT_SPLIT=$S timeout 300 ncu --metrics $M --clock-control none -k regex:gather_kernel -s 3 -c 1 --csv \
    --log-file gpurun_out/gsplit_$S.csv python profiles/ncu_step.py > gpurun_out/gsplit_$S.log 2>&1
  echo "split=$S"; grep rows_gathered gpurun_out/gsplit_$S.log
  grep -o '"[a-z_]*__[a-z_.]*","[A-Za-z%]*","[0-9.,]*"' gpurun_out/gsplit_$S.csv
done
