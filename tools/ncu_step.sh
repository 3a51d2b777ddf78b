timeout 900 ncu --set full --clock-control none --import-source on \
    -k regex:"k_tile_hist|k_aggregate|k_parity|k_pip_cells|k_fused_pure|k_mixed_cells|k_touch" \
    -c 7 -o gpurun_out/full_r01 -f python tools/prof_step.py conus 256 2 four_fused > gpurun_out/full_r01.log 2>&1
