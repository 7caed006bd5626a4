for dbg in 0 2; do ST_DBG=$dbg python tools/quickbench.py 4x256 2>&1 | grep "512 float32 D=3\|256 float32 D=3\|512 float32 D=4"; done
