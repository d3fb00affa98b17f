python -c "import __graft_entry__ as g; g.build()"
python tools/time_filter.py
for v in i16 m3 b8 b2; do NESTGPU_LIB=vlib/$v.so python tools/time_filter.py; done
python tools/time_filter.py
