#!/bin/bash
# final check + profiles in one call
mkdir -p gpurun_out
bash profiles/final_check.sh
bash profiles/round_profile.sh
bash profiles/passb_traffic.sh > gpurun_out/passb_traffic.log 2>&1
ls gpurun_out
