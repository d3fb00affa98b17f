python -c "import __graft_entry__ as g; g.build()"
python tools/time_sort.py
NESTGPU_LIB=vlib/preagg.so python tools/time_sort.py
python tools/time_sort.py
NESTGPU_LIB=vlib/preagg.so python tools/time_sort.py
