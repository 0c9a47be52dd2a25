for L in ${LIBS:-default}; do
  if [ $L = default ]; then export GTR_LIB=$PWD/paper_conf_cgo_hubercgtddcd22_b200/libgtr.so; else export GTR_LIB=$PWD/exp/libgtr_$L.so; fi
  echo "== $L"; python tools/xs_launch.py spmd --time --reps 5 2>&1 | tail -1
  ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct,lts__t_sectors.sum,l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:kernel_rt -c 1 python tools/xs_launch.py spmd 2>&1 | grep -E "dram__|hit_rate|lts__t_sectors|wavefronts|duration"
done
