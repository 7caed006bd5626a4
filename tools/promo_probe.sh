for pr in 0 1 2 3; do echo "promo $pr"; ST_L2PROMO=$pr python tools/quickbench.py 4x256 2>&1 | grep -E "512 float32 D=[34]|256 float32 D=[34]"; done
