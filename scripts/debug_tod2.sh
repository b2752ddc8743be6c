export PYTHONPATH=.
echo "== default"; python scripts/debug_tod.py
echo "== no TMA"; TOASTB200_LIB=vbuild/libtoastb200_notma.so python scripts/debug_tod.py
