ncu --set full --clock-control none --import-source on -k regex:assign_tc -s 1 -c 1 -o gpurun_out/km_epw3 ./scripts/km_prof > /dev/null 2>&1
ls -la gpurun_out/km_epw3*
