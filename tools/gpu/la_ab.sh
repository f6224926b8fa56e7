python tools/la_ab.py c5 lookahead=0,1
python tools/la_ab.py c3 lookahead=0,1
python tools/la_ab.py c4 lookahead=0,1
