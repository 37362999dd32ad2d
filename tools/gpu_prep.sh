for m in 0 1 0 1; do INSTA_PREP_MEMSET=$m timeout 300 python tools/sl_time.py C4 0 0 2>&1 | head -1; done
