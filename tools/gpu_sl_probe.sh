timeout 300 python tools/sl_time.py C3 0 0 2>&1 | grep -E "C3|cone|update"
timeout 300 python tools/sl_time.py C4 0 0 2>&1 | grep -E "C4|cone|update"
