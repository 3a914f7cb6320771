#!/bin/bash
# warm-cache ncu metrics of one PR sweep launch for several vertex orders
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,sm__cycles_active.avg,sm__cycles_active.max,smsp__issue_active.avg.pct_of_peak_sustained_active
for o in ${ORDERS:-none out}; do
  ncu --metrics $M --cache-control none --clock-control none -k regex:${KERN:-k_pr_sell} -s ${SKIP:-8} -c ${COUNT:-1} --csv \
    python tools/relabel_exp.py --scale 24 --orders $o --algos ${ALGOS:-pagerank} --reps 1 > gpurun_out/ncu_relabel_$o.csv 2>&1
done
