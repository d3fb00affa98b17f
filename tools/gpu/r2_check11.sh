python -c "import __graft_entry__ as g; g.build()"
python tools/time_filter.py
NESTGPU_LIB=vlib/i16.so python tools/time_filter.py
NESTGPU_LIB=vlib/i32.so python tools/time_filter.py
