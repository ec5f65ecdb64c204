# GPU: k_sf_gen variants A/B (C4a, C4b) + a full ncu capture of k_sf_gen on C4a (level 3)
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1
VARIANTS="$VARIANTS" CFGS="${CFGS:-C4a C4b}" STEPS=20 bash tools/gpu_variants.sh
if [ -n "$NCU" ]; then KS="$NCU" CFG=C4a S=3 bash tools/gpu_ncu_two.sh; fi
