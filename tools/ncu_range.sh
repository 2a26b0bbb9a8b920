mkdir -p gpurun_out

M=gpu__time_duration.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,dram__bytes_read.sum,dram__bytes_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active,lts__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sectors.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_red.sum,dram__cycles_active.avg.pct_of_peak_sustained_elapsed,fbpa__cycles_active.avg.pct_of_peak_sustained_elapsed
for mode in sample gather full; do
ncu --replay-mode app-range --metrics $M --csv python tools/exp_range_metrics.py --lanes 16 --batches 256 --mode $mode > gpurun_out/range_$mode.csv 2>&1
done
