timeout 600 python tools/cone_cross.py C4
timeout 300 python tools/cone_cross.py C3
