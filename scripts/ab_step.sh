python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for i in 1 2; do
timeout 300 python scripts/diag_step.py 2>&1 | grep -E "pure|hyb_async +f=0.001|hyb_async_allclaims"
DYSEL_LIB=exp_libs/nopdlinit/libdysel.so timeout 300 python scripts/diag_step.py 2>&1 | grep -E "pure|hyb_async +f=0.001"
done
