timeout 200 python profiles/probes/latency_probe.py products
WG_FLAGS=0x20 timeout 200 python profiles/probes/latency_probe.py products
timeout 300 ncu --kernel-name regex:hop_small --launch-count 3 --set full --import-source on -o gpurun_out/hop_small -f python profiles/probes/small_hop_race.py 4 > gpurun_out/ncu_small.log 2>&1
ncu -i gpurun_out/hop_small.ncu-rep --page details --csv > gpurun_out/hop_small_details.csv 2>&1
