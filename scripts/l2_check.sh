cd $GRAFT_REPO_ROOT
for v in 1 0; do
GROPHECY_PF=$v python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1
timeout 600 ncu --metrics lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,dram__bytes_read.sum,gpu__time_duration.sum,lts__t_requests_srcunit_tex.sum --clock-control none -k regex:sweep_kernel -s 3 -c 1 python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline 2>&1 | grep -E "lts__|dram__|gpu__time" 
done
