timeout 600 python exp/rs_variants.py rs-large 0,1,3
