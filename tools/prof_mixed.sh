python tools/mixed_stats.py conus > gpurun_out/mixed_stats.txt 2>&1
for L in default ab/libzh_nogroup.so; do
  if [ "$L" = default ]; then unset ZH_LIBZH; T=grp; else export ZH_LIBZH=$PWD/$L; T=nogrp; fi
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_mixed_cells|k_pip_cells" -c 1 -o gpurun_out/full_$T -f python tools/prof_step.py conus 256 1 fused > gpurun_out/full_$T.log 2>&1
done
