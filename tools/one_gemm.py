import sys, os; sys.path.insert(0,'tools'); sys.path.insert(0,'.')
from gemm_micro import time_linear
M,N,K=map(int,sys.argv[1:4])
print(time_linear(M,N,K,reps=2))
