python -c "import __graft_entry__ as g; g.build()"
python tools/time_filter.py
NESTGPU_LIB=vlib/m6.so python tools/time_filter.py
NESTGPU_LIB=vlib/i4m6.so python tools/time_filter.py
NESTGPU_LIB=vlib/m8.so python tools/time_filter.py
