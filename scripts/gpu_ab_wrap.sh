P=paper_conf_asplos_lucw0cz25_b200
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/memprobe_r01i.csv ./scripts/memprobe > gpurun_out/memprobe_r01i.log 2>&1
./scripts/memprobe > gpurun_out/memprobe_r01i_timed.log 2>&1; cat gpurun_out/memprobe_r01i_timed.log
bash scripts/knob_sweep.sh "BZK_PREFETCH=0" "BZK_PREFETCH=0 BZK_CTA_WAVES=1" "BZK_PREFETCH=0 BZK_CTA_WAVES=2" "BZK_PREFETCH=0 BZK_CTA_WAVES=8" "BZK_PREFETCH=0 BZK_PPT_MAX=16" "BZK_PREFETCH=0 BZK_PPT_MAX=256"
BZK_PREFETCH=0 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    --replay-mode application -k regex:"k_round" -c 11 --csv --log-file gpurun_out/traffic_r01i_nopf.csv \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > /dev/null 2>&1
