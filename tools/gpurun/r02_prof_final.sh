#!/bin/bash
# ncu (application replay) of wc_kernel with the final code, device and host staging, 64 x 16 MiB
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_aperture_sysmem.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,l1tex__throughput.avg.pct_of_peak_sustained_active,sm__throughput.avg.pct_of_peak_sustained_elapsed,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,smsp__inst_executed.sum
python -c "import inputs; inputs.make_corpus(512, 16 << 20)" > /dev/null 2>&1
timeout 900 ncu --replay-mode application --clock-control none --metrics $M -k regex:wc_kernel -c 1 --csv --page raw python tools/prof_wc.py device 64 > $O/r02f_wc_device_ncu_raw.csv 2> $O/r02f_wc_device_ncu.err; echo "wc device ncu rc=$?"
timeout 900 ncu --replay-mode application --clock-control none --metrics $M -k regex:wc_kernel -c 1 --csv --page raw python tools/prof_wc.py host 64 > $O/r02f_wc_host_ncu_raw.csv 2> $O/r02f_wc_host_ncu.err; echo "wc host ncu rc=$?"
