cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/lu_launches.csv python tools/getrf_once.py > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:gemm_syrk -s 8 -c 1 -o gpurun_out/lu_gemm python tools/getrf_once.py > gpurun_out/lu_ncu.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:laswp -s 8 -c 1 -o gpurun_out/lu_laswp python tools/getrf_once.py >> gpurun_out/lu_ncu.log 2>&1
