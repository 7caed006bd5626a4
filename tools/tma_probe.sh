for dbg in 0 1; do ST_DBG=$dbg python tools/quickbench.py "" 2>&1 | grep -E "256 float32 D=[234]|512 float32 D=[34]"; done
