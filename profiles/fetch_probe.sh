#!/bin/bash
# DRAM bytes fetched per gathered row vs row size / L2 fetch granularity (profiles/fetch_probe.py)
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,lts__t_requests_srcunit_tex_op_read.sum
for G in ${GS:-default 32 64}; do
  if [ "$G" = default ]; then unset WG_L2_FETCH; else export WG_L2_FETCH=$G; fi
  timeout 600 ncu --metrics $M --clock-control none -k regex:gather_kernel --csv --log-file gpurun_out/fetch_$G.csv \
      python profiles/fetch_probe.py > gpurun_out/fetch_$G.log 2>&1; echo "$G rc=$?"
done
unset WG_L2_FETCH
python profiles/fetch_table.py gpurun_out/fetch_*.csv
