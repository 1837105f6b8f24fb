LANDAU_LIB=build_variants/liblandau_old.so python scripts/sb_compare.py old_fused
LANDAU_LIB=build_variants/liblandau_old.so LANDAU_FUSED_SINGLE=0 python scripts/sb_compare.py old_multi
python scripts/sb_compare.py new_fused
LANDAU_FUSED_SINGLE=0 python scripts/sb_compare.py new_multi
